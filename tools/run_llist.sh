# ncu launch list (per-kernel durations) of one codec_bench call: $CODEC $MIB $S $DTYPE
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/llist_${CODEC}.csv python tools/codec_bench.py --codecs $CODEC --mib ${MIB:-256} --s ${S:-0.5} --dtype ${DTYPE:-f32} --reps 1 > /dev/null 2>&1
