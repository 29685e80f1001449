# full ncu captures (source-level) of the three step kernels on the E. coli config
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for k in smem_subgraph msp_block scatter_kernel; do
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/p2_$k -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/p2_$k.log 2>&1; echo "$k rc=$?"
done
ls -la gpurun_out
