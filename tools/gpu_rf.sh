cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
python tools/trace_cta.py --config uniform --slot 5 --slot 6
for lib in exp/fc4.so exp/fc3.so exp/fc2.so exp/fc2_cr4.so; do
  ECLMST_LIB=$lib bash tools/gpu_opt_ab.sh "rmat uniform rgg" "-" | sed "s#^#$lib #"
done
