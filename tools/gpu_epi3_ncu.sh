mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/epi3s -f python tools/one_gemm.py 1 3 5376 768 768 0 0 4 > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/epi0s -f python tools/one_gemm.py 1 0 5376 768 768 0 0 4 > /dev/null 2>&1
ls gpurun_out/*.ncu-rep
