#!/bin/bash
# build the library (abort on failure) then run the given command on the GPU box
set -o pipefail
cd /root/repo || exit 1
out=$(timeout 900 python /root/repo/paper_conf_asplos_sivathanucsz19_b200/build.py 2>&1) || { echo "$out" | grep -v warning | tail -20; echo BUILD FAILED; exit 1; }
timeout ${GTO:-2700} /usr/local/graft/bin/gpurun --timeout ${GLIM:-1500} -- "$1" 2>&1 | grep -v "^\[gpurun\] sending"
