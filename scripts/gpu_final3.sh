# Round-1 closing evidence for the current default dispatch: smoke, GPU tests, GPT bench
# (+ torchrun world-1 line, reference arm), ncu launch list, ncu --set full of one pair_step launch.
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 3 --warmup 3 > gpurun_out/bench_gpt.json 2> gpurun_out/bench_gpt.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_gpt_reference.json 2> gpurun_out/bench_gpt_reference.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29531 bench.py --gpus 1 --steps 3 --warmup 3 --no-cpu --force-dist > gpurun_out/bench_gpt_dist.json 2> gpurun_out/bench_gpt_dist.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_gpt.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pair_step -s 200 -c 1 -o gpurun_out/prof_pair_step python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_full.log 2>&1
echo done
