# Build the measurement library libks_dbg.so (never the shipped libks.so): KS_DEBUG work-dropping
# knobs (KS_R1_DEBUG, KS_RV_DEBUG, KS_TC_DEBUG_SKIP_V) and bounded waits, KS_PROF phase clocks,
# KS_TRACE unit timeline.  Select it with KS_LIB=libks_dbg.so.
# Usage: [DEBUG=0|1] [PROF=0|1] [TRACE=0|1] bash tools/build_debug_lib.sh
python -c "
from paper_conf_icppw_wangkbgj16_b200 import build as b
print(b.build_debug(debug=${DEBUG:-1}, prof=${PROF:-1}, trace=${TRACE:-0}))"
