#!/bin/bash
# Build libksel.so of git revision $1 (default HEAD) as paper_conf_ipps_tang0emg15_b200/libksel_A.so
rev=${1:-HEAD}
root=$(cd "$(dirname "$0")/.." && pwd)
rm -rf /tmp/ab_wt && git -C "$root" worktree add -f /tmp/ab_wt "$rev" >/dev/null 2>&1 || exit 1
(cd /tmp/ab_wt && python paper_conf_ipps_tang0emg15_b200/build.py >/dev/null 2>&1) || { echo build failed; exit 1; }
cp /tmp/ab_wt/paper_conf_ipps_tang0emg15_b200/libksel.so "$root/paper_conf_ipps_tang0emg15_b200/libksel_A.so"
git -C "$root" worktree remove --force /tmp/ab_wt
echo "built $rev -> libksel_A.so"
