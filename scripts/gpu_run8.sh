cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/membench tools/membench.cu > gpurun_out/membench_build.log 2>&1
timeout 300 ./tools/membench > gpurun_out/membench.json 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1
timeout 900 python bench.py --config gpt --steps 3 --warmup 3 > gpurun_out/bench_gpt.json 2> gpurun_out/bench_gpt.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_gpt.csv python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_launch.log 2>&1
timeout 900 python scripts/compare_alg1.py --out gpurun_out/alg1_vs_sweep.md > gpurun_out/alg1.log 2>&1
echo done
