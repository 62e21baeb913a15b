mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
K='neighbors_kernel' TAG=nbr_src SKIP=1 COUNT=1 bash tools/ncu_one.sh
K='momentum_energy_kernel' TAG=mom_src SKIP=1 COUNT=1 bash tools/ncu_one.sh
