#!/bin/bash
cd $GRAFT_REPO_ROOT
for f in 0 1 2 6 7; do echo "flags $f"; STRINGS_DISPATCH_FLAGS=$f timeout 120 python tools/latency_probe.py; done
