#!/bin/bash
# local helper: clear gpurun_out/ and run one command on the GPU box (timeout $1 seconds)
cd /root/repo || exit 1
find gpurun_out -mindepth 1 -delete 2>/dev/null
T=$1; shift
exec /usr/local/graft/bin/gpurun --timeout "$T" -- "$@"
