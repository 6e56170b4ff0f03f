for v in tr tailtr; do echo "== trace $v"; CKPT_LIB=variants/lib_$v.so python tools/leaf_trace.py; done
for rep in 1 2; do for v in base tail; do
  echo "== $v"; CKPT_LIB=variants/lib_$v.so python tools/step_timeline.py 20 2>&1 | head -2
done; done
for v in base tail; do echo "== micro $v"; CKPT_LIB=variants/lib_$v.so timeout 300 python tools/leaf_micro.py --gb 3.2 --chunks 4096,512,65536 --modes f32,f64 --reps 20 2>&1 | grep -v "^{"; done
