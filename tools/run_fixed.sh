# fixed per-call cost of the ZVC codec groups: 1 / 4 / 24 MiB, with and without CUDA graphs
for g in 1 0; do for mib in 1 4 24; do
CSWAP_GRAPHS=$g timeout 300 python tools/codec_bench.py --codecs zvc --mib $mib --s 0.5 --reps 20 | python -c "
import sys,json
r=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('graphs $g', r['MiB'], 'MiB c', r['compress']['ms'], 'd', r['decompress']['ms'])"
done; done
