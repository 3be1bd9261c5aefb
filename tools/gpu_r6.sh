mkdir -p gpurun_out
for m in 12 22 2 21; do timeout 120 python tools/probe_modes.py $m 5120 3072 768; done
for m in 12 22; do timeout 120 python tools/probe_modes.py $m 8192 3072 1024; done
for m in 12 22; do timeout 120 python tools/probe_modes.py $m 3072 768 5120 1 1; done
for m in 12 22; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm -s 3 -c 1 -o gpurun_out/mode$m python tools/probe_modes.py $m 5120 3072 768 > gpurun_out/ncu_m$m.log 2>&1
  ncu -i gpurun_out/mode$m.ncu-rep --page raw --csv > gpurun_out/mode${m}_raw.csv 2>/dev/null
  ncu -i gpurun_out/mode$m.ncu-rep --page source --csv --print-source sass > gpurun_out/mode${m}_src.csv 2>/dev/null
done
