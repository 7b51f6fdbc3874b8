# A/B of deferred gather accumulation against the default build.
# The BC_SEQ_PIPE / BC_COOP_PIPE patches were measured slower and removed from
# bc_kernels.cuh; this script is kept as the variant_cmp recipe used for them.
mkdir -p gpurun_out
export VARIANTS="${VARIANTS:-pipe:-DBC_SEQ_PIPE=1}"
SWEEP=tools/gpu/sweep_pipe.txt bash tools/gpu/variant_cmp.sh
