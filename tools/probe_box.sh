nvidia-smi; nvidia-smi topo -m; lscpu | head -30; grep -E "MemTotal|MemAvailable|Hugepage" /proc/meminfo; numactl -H 2>/dev/null | head; df -h /tmp /dev/shm; nproc
python tools/probe_box.py
