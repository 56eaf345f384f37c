timeout 900 python -m pytest tests/test_gpu_graphs.py -x -q -m gpu 2>&1 | tail -2
for cfg in 0 1 3 7 8; do
  echo "== cfg $cfg"
  for d in f32 f16; do for mib in 1024 96; do CSWAP_ZVC_CFG=$cfg timeout 300 python tools/codec_bench.py --codecs zvc --mib $mib --s 0.2,0.5,0.95 --dtype $d 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(r['dtype'], r['MiB'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'])"; done; done
done
