#!/bin/bash
# build locally; only if the build succeeds, run the given command on the GPU box
cd /root/repo
if ! make lib > /tmp/build.log 2>&1; then grep -E "error" /tmp/build.log | head -5; echo "BUILD FAILED"; exit 1; fi
timeout ${TMO:-3000} /usr/local/graft/bin/gpurun --timeout ${GTMO:-1500} -- "$1" 2>&1 | grep -v "^\[gpurun\] sending"
