# K1 CTA shape: interleaved repeats of base vs 4-warp CTAs on the c2 and c5 bench steps
for rep in 1 2 3; do
  bash tools/variant_sweep.sh c2 100
  bash tools/variant_sweep.sh c5 20
done > gpurun_out/cta2.log 2>&1
cat gpurun_out/cta2.log
