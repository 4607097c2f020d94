#!/bin/bash
# Run a command with a host-memory guard: kill it (not the box) if available
# memory drops below GUARD_GB (default 8).  Usage: scripts/run_guarded.sh cmd...
"$@" &
pid=$!
lim=${GUARD_GB:-8}
while kill -0 $pid 2>/dev/null; do
    avail=$(awk '/MemAvailable/{print int($2/1048576)}' /proc/meminfo)
    if [ "$avail" -lt "$lim" ]; then echo "[guard] MemAvailable ${avail} GB < ${lim} GB: killing $pid" >&2; kill -9 $pid; fi
    sleep 1
done
wait $pid
