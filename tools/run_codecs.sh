# parity of the codec kernels + GB/s of RLE / CSR at 256 MiB (iid and clustered)
timeout 900 python -m pytest tests/test_gpu_codecs.py tests/test_gpu_fullsize.py -x -q -m gpu ${PYTEST_K:+-k "$PYTEST_K"} 2>&1 | tail -2
for kind in iid clustered; do for d in f32 f16; do
timeout 300 python tools/codec_bench.py --codecs ${CODECS:-rle,csr} --mib 256 --s 0.5,0.8,0.95 --dtype $d --kind $kind --check 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: r=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print('$kind', r['codec'], r['dtype'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'], 'd', r['decompress']['ms'], r['decompress']['frac'], r.get('roundtrip_ok'))"
done; done
