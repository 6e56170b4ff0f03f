#!/bin/bash
# Co-residency probes: start delay of a PDL-launched 1-warp kernel after the fused leaf kernel,
# for follower bodies of different register counts (variants probe_rNN).
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for v in ${PROBES:-probe_r24 probe_r40 probe_r56 probe_r100}; do
  echo "== $v"
  CKPT_FOLLOW=0 timeout 300 python tools/probe_follow.py variants/$v/libckpt.so
done
