timeout 600 python -m pytest tests/test_gpu_codecs.py -x -q -m gpu -k "lz4 or LZ4" 2>&1 | tail -2
CSWAP_GRAPHS=0 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize.py > gpurun_out/san_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/san_racecheck.log
tail -3 gpurun_out/san_racecheck.log
for d in f32; do timeout 300 python tools/codec_bench.py --codecs lz4 --mib 256 --s 0.5 --kind clustered | cut -c1-220; done
