#!/bin/bash
# scratch driver for one gpurun call: runs the commands given as arguments, logs to gpurun_out/
nproc; free -g | head -2
for c in "$@"; do echo "== $c"; eval "$c"; echo "rc=$?"; done
