mkdir -p gpurun_out
for c in "FFN1 gelu:gf" "FFN2 drop+res:fd" "wgr FFN2 (H:wg"; do
  name="${c%%:*}"; tag="${c##*:}"
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tcp -s 3 -c 1 -o gpurun_out/ncu_$tag python tools/bench_gemm.py 8192 "$name" 1 > gpurun_out/ncu_$tag.log 2>&1; echo "$tag rc=$?"
done
