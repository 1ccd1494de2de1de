set -x
nvidia-smi
nvidia-smi -q | grep -A12 -i "PCI$" | head -40
nvidia-smi -q | grep -iE "Link (Gen|Width)|Current|Max" | head -20
nvidia-smi topo -m
free -g; nproc; lscpu | head -30; numactl -H 2>/dev/null || ls /sys/devices/system/node
cat /proc/meminfo | grep -i huge
ulimit -l
timeout 300 ./tools/probe_link 4096
