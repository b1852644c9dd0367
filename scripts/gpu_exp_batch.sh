cd $GRAFT_REPO_ROOT
timeout 600 python scripts/exp_batch_l2.py gpt 0,64,16,8,4,2 > gpurun_out/exp_batch.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_bytes.sum --clock-control none -k regex:step_persist -s 3000 -c 5 --csv --log-file gpurun_out/exp_ncu_b4.csv python scripts/exp_batch_l2.py gpt 4 > gpurun_out/exp_ncu_b4.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_bytes.sum --clock-control none -k regex:step_persist -s 300 -c 5 --csv --log-file gpurun_out/exp_ncu_b0.csv python scripts/exp_batch_l2.py gpt 0 > gpurun_out/exp_ncu_b0.log 2>&1
echo done
