# per-kernel device durations of 24 / 96 MiB ZVC compress + decompress (ncu launch list, serialised)
for mib in 24 96; do
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/small_$mib.csv python tools/codec_bench.py --codecs zvc --mib $mib --s 0.5 --reps 3 > gpurun_out/small_$mib.log 2>&1
python tools/codec_bench.py --codecs zvc --mib $mib --s 0.5 --reps 20
done
