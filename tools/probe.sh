#!/bin/bash
# Phase-0 box probe: topology, host, link bandwidths. Writes gpurun_out/probe.txt
mkdir -p gpurun_out
{
  echo "== nvidia-smi"; nvidia-smi
  echo "== topo"; nvidia-smi topo -m
  echo "== lscpu"; lscpu
  echo "== nproc"; nproc
  echo "== free"; free -g
  echo "== numactl"; numactl -H 2>&1 || echo "no numactl"
  echo "== ulimit -l"; ulimit -l
  echo "== nvidia-smi -q pcie"; nvidia-smi -q | grep -A12 -i "PCI$\|GPU Link Info\|Link Width\|Max\b" | head -60
  echo "== probe"; timeout 300 ./build/probe ${1:-8}
} > gpurun_out/probe.txt 2>&1
tail -40 gpurun_out/probe.txt
