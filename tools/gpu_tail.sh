for gb in 0.4 0.8 1.6 3.2 6.4 12.8; do
  timeout 300 python tools/leaf_micro.py --gb $gb --chunks 4096 --modes f32 --reps 20 2>&1 | grep -v "^{" | sed "s/^/gb=$gb /"
done
timeout 300 python tools/step_timeline.py > gpurun_out/step_timeline.txt 2>&1
