# usage: bash scratch/launches.sh "<variant>" [tag]
V="$1"; TAG="${2:-cur}"
ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --profile --steps 1 > gpurun_out/p_$TAG.log 2>&1
python profiles/summarise_launches.py gpurun_out/launches_$TAG.csv | head -${3:-12}
