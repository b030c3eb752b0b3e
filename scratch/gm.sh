for gm in 1 4 8 16; do echo "gm=$gm"; ASTRA_GM=$gm python bench_gemm.py --shapes "a1,dU,dX" 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l)
    if d.get('cfg') in ('256.1.1','256.1.1.2','256.1.2'): print('  ', d['shape'][:24].ljust(24), d.get('cfg'), d.get('us'), d.get('tflops'))
"; done
