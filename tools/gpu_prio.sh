for rep in 1 2; do
echo "== lo"; python tools/step_timeline.py 20 2>&1 | head -5
echo "== hi"; CKPT_SIDE_PRIORITY=hi python tools/step_timeline.py 20 2>&1 | head -5
done
