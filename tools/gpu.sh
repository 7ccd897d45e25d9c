#!/bin/bash
# Build locally (abort on failure), then run the given command on the GPU box.
# usage: tools/gpu.sh <timeout_s> '<command>'  (log: /tmp/gpurun_last.log)
set -e
cd /root/repo
python /root/repo/paper_conf_sosp_gonglmc0lwl23_b200/build.py > /tmp/build.log 2>&1 || { tail -20 /tmp/build.log; echo BUILD FAILED; exit 1; }
python -c "import oracle; oracle.build()"
/usr/local/graft/bin/gpurun --timeout "$1" -- "$2"
