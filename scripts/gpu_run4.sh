cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python -m pytest tests -m gpu -q -x -k "toy or fuzz or early or paper or cnn or batch" > gpurun_out/pytest_persist.log 2>&1
timeout 900 python bench.py --config gpt --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_gpt_persist.json 2> gpurun_out/bench_gpt_persist.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:step_persist -s 500 -c 1 -o gpurun_out/prof_persist python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_persist.log 2>&1
echo done
