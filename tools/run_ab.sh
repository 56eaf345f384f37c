timeout 900 python -m pytest tests/test_gpu_codecs.py tests/test_gpu_fullsize.py tests/test_gpu_swap.py -x -q -m gpu 2>&1 | tail -3
for v in "" old vec named; do
  echo "== variant '$v'"
  for d in f32 f16; do CSWAP_LIB_VARIANT=$v timeout 300 python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.2,0.5,0.95 --dtype $d --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(r['dtype'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'], 'd', r['decompress']['ms'], r['decompress']['frac'], r.get('roundtrip_ok'))"; done
done
