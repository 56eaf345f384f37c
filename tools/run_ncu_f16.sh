# ncu --set full with source of the ZVC kernels at 1 GiB: f16 s=0.5 compress, f16 s=0.95, f32 s=0.95
set -x
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:zvc_compress_persistent -s 2 -c 1 -o gpurun_out/f16c_s05 -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.5 --dtype f16 --ncu > gpurun_out/ncu1.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"zvc_(compress_persistent|expand)" -s 4 -c 2 -o gpurun_out/f16_s095 -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.95 --dtype f16 --ncu > gpurun_out/ncu2.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"zvc_(compress_persistent|expand)" -s 4 -c 2 -o gpurun_out/f32_s095 -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.95 --dtype f32 --ncu > gpurun_out/ncu3.log 2>&1
ls -la gpurun_out
