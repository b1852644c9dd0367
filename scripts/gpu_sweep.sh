cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for np_ in 1 2 4; do for tb in 1 8; do
MADPIPE_NPROD=$np_ MADPIPE_TILE_BLOCK=$tb timeout 600 python bench.py --config gpt --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/sweep_${np_}_${tb}.json 2>/dev/null
done; done
echo done
