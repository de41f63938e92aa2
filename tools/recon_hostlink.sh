set -x
mkdir -p gpurun_out
{
lscpu; nproc; cat /proc/meminfo | head -5; which numactl && numactl -H; 
nvidia-smi topo -m; nvidia-smi -q | head -80; 
for d in /sys/bus/pci/devices/*; do if [ "$(cat $d/vendor 2>/dev/null)" = "0x10de" ]; then echo $d numa=$(cat $d/numa_node) speed=$(cat $d/current_link_speed 2>/dev/null) width=$(cat $d/current_link_width 2>/dev/null) class=$(cat $d/class); fi; done
cat /sys/kernel/mm/transparent_hugepage/enabled
ls /sys/class/iommu 2>/dev/null; dmesg 2>/dev/null | grep -i iommu | head
cat /proc/cmdline
} > gpurun_out/recon.txt 2>&1
timeout 600 tools/micro/build/hostlink 32 0 > gpurun_out/hostlink_alloc.txt 2>&1
timeout 600 tools/micro/build/hostlink 32 1 > gpurun_out/hostlink_reg.txt 2>&1
