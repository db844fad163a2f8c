# Build the measurement library libks_dbg.so (never the shipped libks.so): KS_DEBUG work-dropping
# knobs (KS_R1_DEBUG, KS_TC_DEBUG_SKIP_V), KS_PROF phase clocks, KS_TRACE unit timeline.
# Usage: [DEBUG=0|1] [PROF=0|1] [TRACE=0|1] bash tools/build_debug_lib.sh
KS_EXTRA_NVCC="-DKS_DEBUG=${DEBUG:-1} -DKS_PROF=${PROF:-1} -DKS_TRACE=${TRACE:-0}" python -c "
from paper_conf_icppw_wangkbgj16_b200 import build as b
b.BUILD=b.BUILD+'_dbg'; b.LIB=b.LIB.replace('libks.so','libks_dbg.so')
print(b.build())"
