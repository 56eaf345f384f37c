timeout 900 python -m pytest tests/test_gpu_codecs.py tests/test_gpu_fullsize.py tests/test_gpu_graphs.py -x -q -m gpu 2>&1 | tail -2
for d in f16 bf16; do for mib in 1024 96; do timeout 300 python tools/codec_bench.py --codecs zvc --mib $mib --s 0.0,0.2,0.5,0.8,0.95 --dtype $d --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(r['dtype'], r['MiB'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'], 'd', r['decompress']['frac'], r.get('roundtrip_ok'))"; done; done
