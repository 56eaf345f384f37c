set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -15 > gpurun_out/s3_pytest.log
timeout 600 python bench.py > gpurun_out/s3_bench.log 2>&1
for d in f32 f16 bf16; do timeout 300 python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.2,0.5,0.8,0.95 --dtype $d; done > gpurun_out/s3_zvc.log 2>&1
timeout 600 python tools/codec_bench.py --codecs rle,csr,lz4 --mib 256 --s 0.5,0.8 > gpurun_out/s3_other.log 2>&1
tail -3 gpurun_out/s3_pytest.log; tail -c 3000 gpurun_out/s3_bench.log
