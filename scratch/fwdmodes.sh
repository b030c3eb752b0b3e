for v in "fwd=0" "fwd=1" "fwd=2"; do
  ASTRA_VARIANT="$v" python bench.py --profile --steps 3 2>&1 | tail -1 | python -c "import sys,json; d=json.loads(sys.stdin.read()); print('$v', {k: round(v,3) for k,v in d['regions_ms'].items()})"
done
ASTRA_VARIANT="fwd=2" ncu --set full --clock-control none --cache-control none --import-source on --kernel-name-base demangled -k regex:"lstm_rec_fwd" -c 1 -o gpurun_out/recfwd_full python bench.py --profile --steps 1 > /dev/null 2>&1
ls gpurun_out/*.ncu-rep
