#!/bin/bash
# generic GPU-box runner: build, then the commands given as arguments (each a
# quoted shell line), outputs under gpurun_out/
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.txt 2>&1 || { echo "build failed"; tail gpurun_out/build.txt; exit 1; }
for c in "$@"; do echo "== $c"; bash -c "$c"; echo "rc=$?"; done
