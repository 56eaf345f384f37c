R=/tmp/ncu_reps; mkdir -p $R
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"lz4_(compress|decode)_kernel" -s 2 -c 4 -o $R/lz4 -f python tools/codec_bench.py --codecs lz4 --mib 4 --s 0.5 --ncu > gpurun_out/ncu_lz4.log 2>&1
python tools/ncu_lines.py $R/lz4.ncu-rep lz4_decode 30 > gpurun_out/lines_lz4_decode.txt 2>&1
python tools/ncu_lines.py $R/lz4.ncu-rep lz4_compress 30 > gpurun_out/lines_lz4_compress.txt 2>&1
ncu -i $R/lz4.ncu-rep --page raw --csv > gpurun_out/raw_lz4.csv 2>&1
