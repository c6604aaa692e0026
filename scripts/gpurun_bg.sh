#!/bin/bash
# usage: scripts/gpurun_bg.sh LOGFILE 'command...'   (runs gpurun in the background from the repo root)
cd /root/repo || exit 1
python -c "import __graft_entry__ as g; g.build()" || exit 1
LOG=$1; shift
( timeout 3000 /usr/local/graft/bin/gpurun --timeout 2400 -- "$@" > "$LOG" 2>&1; echo EXIT $? >> "$LOG" ) > /dev/null 2>&1 &
echo "started -> $LOG"
