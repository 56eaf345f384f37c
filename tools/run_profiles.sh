# Round-end evidence with the current kernels: GPU tests, bench line, ncu launch list of the bench
# command, ncu --set full summaries of the bench step's compress / decode launches and of the
# 1 GiB micro kernels.  Outputs in gpurun_out/ (copied to profiles/ by hand).
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks_throttle_reasons.active --format=csv
timeout 1500 python -m pytest tests -q -m gpu -x 2>&1 | tail -3 > gpurun_out/p_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/p_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/p_smoke.log
timeout 900 python bench.py > gpurun_out/p_bench.json 2> gpurun_out/p_bench.err
timeout 900 python bench.py --workload bert --no-cpu > gpurun_out/p_bench_bert.json 2> gpurun_out/p_bench_bert.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/p_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/p_launches.log 2>&1
timeout 1200 ncu --set full --clock-control none -k regex:zvc_compress -s 36 -c 12 -o gpurun_out/p_bench_step -f python bench.py --steps 1 --warmup 3 --no-extras --no-cpu > gpurun_out/p_ncu1.log 2>&1
timeout 1200 ncu --set full --clock-control none -k regex:"zvc_(count|scan|expand)" -s 378 -c 30 -o gpurun_out/p_bench_dec -f python bench.py --steps 1 --warmup 3 --no-extras --no-cpu > gpurun_out/p_ncu2.log 2>&1
for d in f32 f16; do
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"zvc_(compress_persistent|expand)" -s 2 -c 2 -o gpurun_out/p_micro_$d -f python tools/codec_bench.py --codecs zvc --mib 1024 --s 0.5 --dtype $d --ncu > gpurun_out/p_ncu_micro_$d.log 2>&1
done
sync; ls -la gpurun_out
