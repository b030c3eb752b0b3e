# usage: bash scratch/ab_lib.sh BASE_SO [reps]   — A/B of the cfg5 step: BASE_SO vs the in-tree build
for i in $(seq ${2:-2}); do
  ASTRA_LIB_OVERRIDE=$1 AB_TAG=base python scratch/ab.py 8 2>&1 | tail -1
  AB_TAG=new python scratch/ab.py 8 2>&1 | tail -1
done
