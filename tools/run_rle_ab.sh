for v in "" $VARIANTS; do echo "== '$v'"; for kind in iid clustered; do
CSWAP_LIB_VARIANT=$v timeout 300 python tools/codec_bench.py --codecs ${CODECS:-rle} --mib 256 --s 0.5,0.95 --kind $kind --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print('$kind', r['codec'], r['dtype'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'], 'd', r['decompress']['ms'], r['decompress']['frac'], r.get('roundtrip_ok'))"
done; done
