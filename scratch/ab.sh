# usage: bash scratch/ab.sh "ENV_A" "ENV_B" [reps]
for i in $(seq ${3:-2}); do
  for cfg in "$1" "$2"; do env $cfg AB_TAG="$cfg" python scratch/ab.py 8 2>&1 | tail -1; done
done
