# Round-end evidence with the current kernels: GPU tests, smoke, bench lines, ncu launch list of
# the bench command, ncu --set full summaries (bench step compress / decode launches, 1 GiB
# micro kernels).  Large .ncu-rep files are summarised on the box and deleted (gpurun copies
# back at most 64 MiB of gpurun_out/).
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_throttle_reasons.active --format=csv
timeout 1500 python -m pytest tests -q -m gpu -x 2>&1 | tail -3 > gpurun_out/p_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/p_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/p_smoke.log
timeout 900 python bench.py > gpurun_out/p_bench.json 2> gpurun_out/p_bench.err
timeout 900 python bench.py --workload bert --no-cpu > gpurun_out/p_bench_bert.json 2> gpurun_out/p_bench_bert.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/p_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/p_launches.log 2>&1
python tools/launch_summary.py gpurun_out/p_launches.csv "python bench.py --steps 2 --warmup 3 --no-extras --no-cpu (under ncu; 5 steps of the VGG16 b64 set incl. warm-up, then the isolated replay of the 12 tensors x 4)" > gpurun_out/p_launches.txt
R=/tmp/ncu_reps; mkdir -p $R
timeout 1200 ncu --set full --clock-control none -k regex:zvc_compress -s 36 -c 12 -o $R/bench_step -f python bench.py --steps 1 --warmup 3 --no-extras --no-cpu > gpurun_out/p_ncu1.log 2>&1
timeout 1200 ncu --set full --clock-control none -k regex:"zvc_(count|scan|expand)" -s 378 -c 30 -o $R/bench_dec -f python bench.py --steps 1 --warmup 3 --no-extras --no-cpu > gpurun_out/p_ncu2.log 2>&1
for d in f32 f16; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"zvc_(compress_persistent|expand)" -s 2 -c 2 -o $R/micro_$d -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.5 --dtype $d --ncu > gpurun_out/p_ncu_micro_$d.log 2>&1
python tools/ncu_sass_mix.py $R/micro_$d.ncu-rep zvc_compress 25 > gpurun_out/p_sassmix_compress_$d.txt 2>&1
python tools/ncu_lines.py $R/micro_$d.ncu-rep zvc_compress 40 > gpurun_out/p_lines_compress_$d.txt 2>&1
done
python tools/ncu_summary.py gpurun_out/p_ncu.json bench_step=$R/bench_step.ncu-rep bench_step_dec=$R/bench_dec.ncu-rep micro_1GiB_f32_s05=$R/micro_f32.ncu-rep micro_1GiB_f16_s05=$R/micro_f16.ncu-rep > /dev/null
cp $R/micro_f16.ncu-rep gpurun_out/p_micro_f16.ncu-rep
sync; ls -la gpurun_out; du -sh gpurun_out
