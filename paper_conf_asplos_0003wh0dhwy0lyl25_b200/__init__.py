"""B200-native TempGraph: chain-driven temporal path queries (EAT, LD, fastest,
shortest, reachability) behind the C-ABI of include/tg.h.

    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import Graph
    g = Graph(n, u, v, t, dur).build()
    arrival = g.query("eat", sources=[0, 5], window=(0, 1000))
"""
from .tempgraph import (  # noqa: F401
    PROBLEMS, TG_EAT, TG_FASTEST, TG_LD, TG_REACH, TG_SHORTEST, TG_TMAX, TG_UNREACHED, Graph, TGError,
    as_u32, load_library, tg_build_chains, tg_export_chains, tg_graph_create, tg_graph_destroy, tg_graph_info,
    tg_kernel_launch_count, tg_last_query_stats, tg_nccl_unique_id, tg_comm_create, tg_comm_destroy,
    tg_graph_attach_comm, tg_profile_enable, tg_query_topk, tg_query_summary, TG_LD_SOURCE, tg_graph_insert_edges, tg_profile_report, tg_release_cached_memory, tg_query, tg_set_option,
)
