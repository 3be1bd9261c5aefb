# In-step CUPTI timeline (tools/trace_step.py) + the per-shape GEMM tile sweep.
mkdir -p gpurun_out/trace
timeout 600 python tools/trace_step.py bert-base 10 gpurun_out/trace/bb.json > gpurun_out/trace/bb.txt 2>&1; echo "trace rc=$?"; cat gpurun_out/trace/bb.txt
MIMOSE_GROUPED_SPLIT=0 timeout 600 python tools/trace_step.py bert-base 10 /tmp/bb0.json > gpurun_out/trace/bb_nosplit.txt 2>&1; echo "trace0 rc=$?"; head -60 gpurun_out/trace/bb_nosplit.txt
gzip -f gpurun_out/trace/bb.json
bash tools/gpu_tile_sweep.sh
