// omprt -- B200-native OpenMP device runtime for offloaded `target teams distribute
// parallel for` (Doerfert et al., IPDPS'22, §III), header-only, compiled into each kernel's
// translation unit -- the analog of linking the runtime bitcode into the application and
// optimizing them together (§II-B).
//
// Device API:
//   Team<Tr> init<Tr>()                                   P:100-112  state.cuh
//   deinit<Tr, Regions, LastWasTerminal>(team)            P:92       parallel.cuh
//   distribute_parallel_for(team, n, body)                Fig. 5     workshare.cuh
//   distribute(team, n, body), for_static(team, n, body)  Fig. 5/Q2  workshare.cuh
//   parallel<Tr, Regions, R>(team, args, num_threads)     P:92       parallel.cuh
//   worker_state_machine<Tr, Regions>(team)               P:92       parallel.cuh
//   alloc_shared(team, bytes), free_shared(team, p, bytes) P:110-112 stack.cuh
//   team_reduce / team_reduce_to_main / league_reduce     north_star reduction.cuh
//   get_thread_num / get_num_threads / get_level / ...    P:102-108  icv.cuh
//   aligned_barrier(), conditional_write()                Fig. 6/7b  sync.cuh
#pragma once
#include "config.cuh"
#include "env.cuh"
#include "icv.cuh"
#include "parallel.cuh"
#include "reduction.cuh"
#include "stack.cuh"
#include "state.cuh"
#include "sync.cuh"
#include "workshare.cuh"
