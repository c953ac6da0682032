mkdir -p gpurun_out/dd2
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sshopm_dedup -s 3 -c 1 -o gpurun_out/dd2/prof_dedup python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/dd2/ncu.log 2>&1
