timeout 900 python -m pytest tests/test_gpu_codecs.py tests/test_gpu_fullsize.py tests/test_gpu_swap.py tests/test_gpu_swap_more.py tests/test_gpu_graphs.py -x -q -m gpu 2>&1 | tail -2
for m in 1 24 96 1024; do for d in f32 f16; do timeout 300 python tools/codec_bench.py --codecs zvc --mib $m --s 0.5 --dtype $d --check | python -c "
import sys,json
r=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(r['dtype'], r['MiB'], 'c', r['compress']['ms'], 'd', r['decompress']['ms'], r['decompress']['frac'], r.get('roundtrip_ok'))"; done; done
