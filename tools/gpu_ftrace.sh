#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
timeout 300 python tools/probe_follow.py variants/ftrace/libckpt.so --ftrace
timeout 600 python tools/probe_follow.py variants/ftrace/libckpt.so --ftrace --c5
