#!/bin/bash
# Build the package of another commit into ab_<name>/ for same-session A/B
# timing (tools/knob_sweep.py with GALLATIN_PKG_ROOT=$PWD/ab_<name>).
# Usage: tools/ab_build.sh <commit> <name>.  ab_*/ is scratch (git-ignored).
set -e
rm -rf /tmp/ab_wt_$2 ab_$2
git worktree add -q /tmp/ab_wt_$2 $1
(cd /tmp/ab_wt_$2 && python -c "
import importlib.util
s = importlib.util.spec_from_file_location('b', 'paper_conf_ppopp_mccoyp24_b200/build.py')
b = importlib.util.module_from_spec(s); s.loader.exec_module(b); b.build()" > /dev/null)
mkdir -p ab_$2 && cp -r /tmp/ab_wt_$2/paper_conf_ppopp_mccoyp24_b200 ab_$2/
git worktree remove --force /tmp/ab_wt_$2
echo "built $1 into ab_$2"
