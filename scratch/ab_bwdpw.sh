# A/B: backward pointwise kernel, cp.async double-buffered rows (default) vs register loads (ASTRA_BWD_PW=0)
rm -f gpurun_out/ab_summary.txt
run() {
  timeout 300 env $1 python bench.py > gpurun_out/ab.log 2>&1
  echo "$1 $(python scratch/ab_summ.py gpurun_out/ab.log 2>&1 | tail -1)" >> gpurun_out/ab_summary.txt
}
for rep in 1 2; do
  for s in "ASTRA_BWD_PW=0" "ASTRA_BWD_PW=1"; do run "$s"; done
done
cat gpurun_out/ab_summary.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lstm_bwd_pw -s 150 -c 1 -o gpurun_out/s4_bwdpw_async python bench.py --profile --steps 1 > /dev/null 2>&1
