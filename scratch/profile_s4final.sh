# Round-1 session-4 profile pass: bench line + launch list of one tuned cfg5 step.  Writes gpurun_out/s4final_*.
python bench.py > gpurun_out/s4final_bench.log 2>&1
V=$(tail -1 gpurun_out/s4final_bench.log | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V" > gpurun_out/s4final_variant.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/s4final_launches_cfg5_step.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/s4final_launches_cfg5_step.csv > gpurun_out/s4final_launches_summary.txt
python bench_micro.py --json gpurun_out/s4final_micro.json > /dev/null 2>&1
tail -1 gpurun_out/s4final_bench.log | cut -c1-400; head -8 gpurun_out/s4final_launches_summary.txt
