V="a1=256.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.2,head=256.1.1.2,wg_side=1,fwd=0,bwd=0"
for m in x; do
ASTRA_BWD_PW=$m ASTRA_VARIANT="$V" python bench.py --profile --steps 5 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$m', {k: round(v,3) for k,v in d['regions_ms'].items()})"
done
ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none -k regex:"lstm_bwd_pw" -s 100 -c 20 --csv --log-file gpurun_out/ab.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/ab.csv | head -3
