# DESIGN §6.1 table: ZVC compress / decompress, 1 GiB x f32 / f16 / bf16 x s, and 96 / 24 MiB f32
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
{ for d in f32 f16 bf16; do timeout 300 python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.2,0.5,0.8,0.95 --dtype $d --check; done
  timeout 300 python tools/codec_bench.py --codecs zvc --mib 96 --s 0.5 --check
  timeout 300 python tools/codec_bench.py --codecs zvc --mib 24 --s 0.5 --check; } > gpurun_out/zvc_table.jsonl 2>&1
python -c "
import json
for l in open('gpurun_out/zvc_table.jsonl'):
    try: r=json.loads(l)
    except Exception: continue
    print(r['dtype'], r['MiB'], r['s'], 'c', r['compress']['ms'], r['compress']['frac'], 'dc', r['decompress']['ms'], r['decompress']['frac'], r.get('roundtrip_ok'))"
