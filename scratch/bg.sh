python bench_gemm.py --shapes "${1:-per step}" 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d['shape'][:44].ljust(44), d.get('cfg'), d.get('us'), d.get('tflops'), d.get('error',''))
"
