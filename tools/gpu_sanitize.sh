# compute-sanitizer over one small step: memcheck on both paths, racecheck and synccheck
mkdir -p gpurun_out/san
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 900 $CS --tool memcheck --leak-check full python tools/sanitize_step.py both > gpurun_out/san/memcheck.log 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/san/memcheck.log
timeout 900 $CS --tool racecheck python tools/sanitize_step.py both > gpurun_out/san/racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/san/racecheck.log
timeout 900 $CS --tool synccheck python tools/sanitize_step.py both > gpurun_out/san/synccheck.log 2>&1; echo "synccheck rc=$?"; tail -3 gpurun_out/san/synccheck.log
timeout 900 $CS --tool initcheck python tools/sanitize_step.py toy > gpurun_out/san/initcheck.log 2>&1; echo "initcheck rc=$?"; tail -3 gpurun_out/san/initcheck.log
