OUT=gpurun_out/sanitize_r02d SIZES="10" bash tools/sanitize.sh
tail -3 gpurun_out/sanitize_r02d/memcheck.log; tail -3 gpurun_out/sanitize_r02d/racecheck.log; tail -3 gpurun_out/sanitize_r02d/synccheck.log
