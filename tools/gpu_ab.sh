# A/B of variants/lib_*.so on the bench step: usage bash tools/gpu_ab.sh "v1 v2" [reps]
for rep in $(seq ${2:-2}); do for v in $1; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so python tools/step_timeline.py 10 2>&1 | head -5
done; done
