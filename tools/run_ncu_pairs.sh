for v in pairs ""; do
CSWAP_LIB_VARIANT=$v ncu --set full --import-source on --clock-control none -k regex:zvc_compress_persistent -s 2 -c 1 -o gpurun_out/c16_$v -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.5 --dtype f16 --ncu > gpurun_out/ncu_c16_$v.log 2>&1
done
sync
