# A/B of the chain GEMMs' shared-memory caps (co-residency of the pointwise kernels), interleaved;
# one line per setting in gpurun_out/ab_summary.txt
run() {
  timeout 300 env $1 python bench.py > gpurun_out/ab.log 2>&1
  echo "$1 $(python scratch/ab_summ.py gpurun_out/ab.log 2>&1 | tail -1)" >> gpurun_out/ab_summary.txt
}
for rep in 1 2; do
  for s in "ASTRA_X=0" "ASTRA_BPTT_SMEM_KB=176" "ASTRA_BPTT_SMEM_KB=176 ASTRA_REC_SMEM_KB=144"; do run "$s"; done
done
cat gpurun_out/ab_summary.txt
