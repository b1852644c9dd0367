cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1
timeout 900 python bench.py --config gpt --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_gpt.json 2> gpurun_out/bench_gpt.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:trans_kernel -s 500 -c 1 -o gpurun_out/prof_trans python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_trans.log 2>&1
echo done
