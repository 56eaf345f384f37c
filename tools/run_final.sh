# Round-end check with the final tree: GPU tests, smoke, bench lines (VGG16 default, ResNet-50,
# BERT), the torchrun launch path (1 process; NCCL max-over-ranks) and the reference arm.
set -x
timeout 1500 python -m pytest tests -q -m gpu 2>&1 | tail -3 > gpurun_out/f_pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/f_smoke.log
timeout 900 python bench.py > gpurun_out/f_bench.json 2> gpurun_out/f_bench.err
timeout 900 python bench.py --workload resnet50 --no-cpu > gpurun_out/f_bench_resnet.json 2> gpurun_out/f_bench_resnet.err
timeout 900 python bench.py --workload bert --no-cpu > gpurun_out/f_bench_bert.json 2> gpurun_out/f_bench_bert.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 1 --steps 3 --warmup 3 --no-extras --no-cpu > gpurun_out/f_torchrun.json 2> gpurun_out/f_torchrun.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/f_ref.json 2> gpurun_out/f_ref.err
