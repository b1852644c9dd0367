# Pair-path GPU tests, then the GPT bench (and the batch bench if BATCH=1) on the current build.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi.py -x -q > gpurun_out/ck_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/ck_pytest.log
tail -3 gpurun_out/ck_pytest.log
for i in 1 2; do timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/ck_gpt_$i.json 2> gpurun_out/ck_gpt_$i.err; done
if [ "${BATCH:-0}" = 1 ]; then timeout 900 python bench.py --config batch --steps 3 --warmup 3 --no-cpu --no-e2e > gpurun_out/ck_batch.json 2> gpurun_out/ck_batch.err; fi
echo done
