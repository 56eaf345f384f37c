for d in f32 f16; do
CSWAP_LIB_VARIANT=named ncu --set full --import-source on --clock-control none -k regex:zvc_compress_persistent -s 2 -c 1 -o gpurun_out/named_$d -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.5 --dtype $d --ncu > gpurun_out/ncu_named_$d.log 2>&1
done
sync; ls -la gpurun_out
