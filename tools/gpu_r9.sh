mkdir -p gpurun_out
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:k_gemm_tc --csv --log-file gpurun_out/gemm_dram.csv python bench.py --steps 3 --warmup 3 --no-baselines --no-cpu-baseline > gpurun_out/ncu_dram.log 2>&1; echo "dram rc=$?"
python tools/gemm_traffic.py gpurun_out/gemm_dram.csv gpurun_out/gemm_traffic.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file gpurun_out/launches_rl.csv python bench.py --config roberta-large --steps 2 --warmup 1 --no-cpu-baseline --no-baselines > gpurun_out/ncu_rl.log 2>&1; echo "rl rc=$?"
python profiles/summarize_launches.py gpurun_out/launches_rl.csv | head -20
