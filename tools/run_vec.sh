set -x
timeout 900 python -m pytest tests/test_gpu_codecs.py tests/test_gpu_fullsize.py -x -q -m gpu 2>&1 | tail -3
for d in f32 f16; do timeout 300 python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.0,0.2,0.5,0.8,0.95 --dtype $d --check; done 2>&1 | cut -c1-260
timeout 300 python tools/codec_bench.py --codecs zvc --mib 96 --s 0.5 --dtype f32 | cut -c1-260
ncu --set full --import-source on --clock-control none -k regex:zvc_compress_persistent -s 2 -c 1 -o gpurun_out/f16c_vec -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.5 --dtype f16 --ncu > gpurun_out/ncu_vec.log 2>&1
sync; ls -la gpurun_out/
