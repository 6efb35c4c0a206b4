#!/bin/bash
# build locally (fail fast), then run the given command on the B200 box
set -e
cd /root/repo
python paper_conf_ipps_fallinadcb25_b200/_build.py > /tmp/build.log 2>&1 || { grep -E "error" /tmp/build.log | head; echo BUILD FAILED; exit 1; }
/usr/local/graft/bin/gpurun --timeout "${GPU_TIMEOUT:-1500}" -- "$@"
