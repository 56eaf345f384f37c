for v in "" b32 b8 u4 sl4; do echo "== variant '$v'"
for d in f32 f16; do for mib in 1024; do CSWAP_LIB_VARIANT=$v timeout 300 python tools/codec_bench.py --codecs zvc --mib $mib --s 0.2,0.5,0.95 --dtype $d --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(r['dtype'], r['MiB'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'], r.get('roundtrip_ok'))"; done; done; done
