# ncu --set full (with source) of the GELU and dropout-residual epilogue GEMMs
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/epi2 -f python tools/one_gemm.py 1 2 5376 3072 768 0 0 4 > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/epi3 -f python tools/one_gemm.py 1 3 5376 768 3072 0 0 4 > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/epi0 -f python tools/one_gemm.py 1 0 5376 3072 768 0 0 4 > /dev/null 2>&1
ls gpurun_out/*.ncu-rep
