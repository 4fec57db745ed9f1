# NUMA placement of the pinned host arrays vs zero-copy gather rate
nvidia-smi topo -m 2>&1 | head -8
lscpu | grep -iE "numa|^CPU\(s\)|Model name"
cat /sys/bus/pci/devices/0000:$(nvidia-smi --query-gpu=pci.bus_id --format=csv,noheader | cut -d: -f2-3 | tr 'A-F' 'a-f')/numa_node 2>/dev/null
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/zc_align tools/zc_align.cu
for n in $(ls -d /sys/devices/system/node/node* | sed 's/.*node//'); do
  cpus=$(cat /sys/devices/system/node/node$n/cpulist)
  echo "== node $n cpus $cpus"
  taskset -c $cpus timeout 300 /tmp/zc_align | grep -E "L=  1024 (16B ld|8B ld)|L= 65536 16B ld" | grep "grid=148"
done
