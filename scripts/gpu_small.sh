cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in resnet50 vgg19 inception_v3; do
  for k in persist v1 tma; do
    MADPIPE_KERNEL=$k timeout 600 python bench.py --config $c --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/small_${c}_${k}.json 2>/dev/null
  done
done
echo done
