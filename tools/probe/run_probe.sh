set -x
mkdir -p gpurun_out
nvidia-smi -L > gpurun_out/box_facts.txt 2>&1
nvidia-smi topo -m >> gpurun_out/box_facts.txt 2>&1
nvidia-smi -q | grep -iE 'pcie|link|gen|width' | head -40 >> gpurun_out/box_facts.txt 2>&1
lscpu >> gpurun_out/box_facts.txt 2>&1
nproc >> gpurun_out/box_facts.txt
free -g >> gpurun_out/box_facts.txt
timeout 300 ./tools/probe/host_link_probe $((1<<30)) > gpurun_out/host_link_probe.json 2> gpurun_out/host_link_probe.err
cat gpurun_out/host_link_probe.json
