cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q -k "toy or fuzz or early or paper" > gpurun_out/pytest_small.log 2>&1
timeout 600 python bench.py --config resnet50 --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_resnet.json 2> gpurun_out/bench_resnet.err
timeout 900 python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/bench_gpt.json 2> gpurun_out/bench_gpt.err
echo done
