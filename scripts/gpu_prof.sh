cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
MADPIPE_PROF=1 timeout 600 python bench.py --config gpt --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/bench_prof.json 2> gpurun_out/bench_prof.err
echo done
