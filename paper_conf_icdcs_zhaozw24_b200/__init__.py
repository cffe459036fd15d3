"""B200-native AdapCC hot path: strategy-driven AllReduce / AllGather / AlltoAll
with ready-mask partial aggregation and relays (§IV-C, §IV-D, §V).

The engine is libadapcc.so (C ABI, include/adapcc.h); ``adapcc`` is the thin
ctypes binding and ``generator`` emits strategy text.
"""

from . import coordinator, costmodel, ddp, generator  # noqa: F401
from .adapcc import (AdapccError, Communicator, plan_items, plan_stats, strategy_check,  # noqa: F401
                     strategy_partition, strategy_sub, strategy_tuples, lib_path)
