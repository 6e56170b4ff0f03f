for v in ${1:-base lvsmall}; do echo "== $v"; CKPT_LIB=variants/lib_$v.so python tools/levels_micro.py; CKPT_LIB=variants/lib_$v.so python tools/step_timeline.py | head -5; done
