#!/bin/bash
# records path: variant builds (steps per trip) x refill K on C2
mkdir -p gpurun_out
for lib in ${LIBS:-variants/rec2.so variants/rec3.so}; do
  SSHOPM_LIBRARY=$PWD/$lib python tools/rec_sweep.py --config ${CFG:-C2} --sets "${SETS:-4:32,2:32,8:32}" --reps 5 2>&1 | grep -v warn | sed "s#^#$(basename $lib) #" | tee -a gpurun_out/rec_var.txt
done
