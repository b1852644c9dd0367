cd $GRAFT_REPO_ROOT
timeout 300 ./tools/tmarate > gpurun_out/tmarate.jsonl 2>&1
