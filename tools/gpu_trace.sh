#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
for d in 0 22; do echo "== HIOS_DBG=$d"; HIOS_DBG=$d timeout 300 python tools/conv_trace.py stem2a 4a 2>&1 | tail -40; done
