# A/B of the persistent ZVC compress: default build vs variant builds (tools/build_variants.py,
# VARIANTS="tag ...") and launch variants (CFGS="0 9 ...", CSWAP_ZVC_CFG)
timeout 900 python -m pytest tests/test_gpu_codecs.py tests/test_gpu_graphs.py -x -q -m gpu 2>&1 | tail -2
for v in "" $VARIANTS; do for cfg in ${CFGS:-0}; do echo "== variant '$v' cfg $cfg"
for d in f32 f16; do CSWAP_ZVC_CFG=$cfg CSWAP_LIB_VARIANT=$v timeout 300 python tools/codec_bench.py --codecs zvc --mib ${MIB:-1024} --s 0.2,0.5,0.95 --dtype $d --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(r['dtype'], r['MiB'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'], r.get('roundtrip_ok'))"; done; done; done
