"""B200 (sm_100a) Bitwise Parallel Bulk Computation of the Smith-Waterman
algorithm (Nishimura, Bordim, Ito, Nakano, IPDPSW 2017).

Public API (same names as the C ABI in include/bpbc_sw.h):
  score_batch, score_batch_host, pack, untranspose, workspace_bytes,
  get_error_flags, last_plan; multi-GPU: parallel.score_sharded.
"""
from ._lib import BPBCError, LIB_PATH  # noqa: F401
from .api import (check_flags, default_score_bits, destroy_all, filter_batch,  # noqa: F401
                  get_error_flags, last_plan, pack, profile, profile_read, release_thread_ctx,
                  score_batch, score_batch_host, score_batch_host_packed2, score_batch_packed2,
                  score_batch_wordwise, untranspose, workspace_bytes, workspace_bytes_for)
from .parallel import (gather_scores, score_multi_device, score_sharded, shard_range,  # noqa: F401
                       shard_ranges)
