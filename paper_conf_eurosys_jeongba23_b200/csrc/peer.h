// Multi-process parallel transmission (one process per GPU): the NCCL send/recv gather.
#pragma once
#include <vector>

#include "engine.h"

namespace dp {

// Slot s of a plan is served by the rank dp_peer_set_slot_ranks named for this primary, else by
// rank (primary + s) % nranks.
int peer_rank_of_slot(const dp_context* ctx, int primary, int slot);

// Primary: post the receives of every PT slot into the model's HBM slots, one NCCL group
// per round (piece r of every secondary), one event per round bound to its units.
void peer_recv_all(dp_context* ctx, dp_model* m, const dp_plan* plan, int prim_rank, int dev, cudaEvent_t fork,
                   std::vector<cudaEvent_t>& unit_ev, dp_run_stats& st);
// Primary: make `exec` wait for every posted receive.
void peer_join(dp_context* ctx, cudaStream_t exec);
// Secondary rank: H2D its slot's pieces into the staging ring and send them to the primary.
void peer_send_rank(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, dp_run_stats* stats);
void peer_destroy(dp_context* ctx);

// The piece list of one slot (shared by sender and receiver so both sides agree).
std::vector<Piece> slot_pieces(const dp_model* m, const dp_plan* plan, int slot, int64_t cap, int64_t tail);
inline int64_t opt_cap(const dp_context* ctx) { return ctx->opts.chunk_bytes < 4096 ? 4096 : ctx->opts.chunk_bytes; }
inline int64_t opt_tail(const dp_context* ctx) { return ctx->opts.tail_bytes; }
void bind_units(std::vector<cudaEvent_t>& unit_ev, const Piece& p, cudaEvent_t e);

// SM-driven forwarder (pt_forward.cu).  go/counter/done are null in one process.
void launch_pt_forward(const void* src, void* dst, int64_t bytes, cudaStream_t s, const uint32_t* go,
                       uint32_t epoch, uint32_t* counter, uint32_t* done);
// Across processes (CUDA IPC mailboxes): the primary releases `go` to its secondaries, then
// waits on done[slot][piece] before the units of that piece; a secondary forwards its slot.
void launch_pt_wait(const uint32_t* flag, uint32_t value, cudaStream_t s);  // one-thread acquire-spin
void ipc_check_primary(dp_context* ctx);
// The primary's kernels read the epoch from its mailbox word, set (outside any graph) by
// ipc_set_epoch before each cold start, so a captured cold-start graph is replayable.
void ipc_set_epoch(dp_context* ctx, uint32_t epoch, cudaStream_t exec);
void ipc_primary_begin(dp_context* ctx, const dp_plan* plan, int prim_rank, cudaStream_t exec);
void ipc_primary_wait(dp_context* ctx, int slot, size_t piece, cudaStream_t exec);
// One wait kernel for several (slot, piece) done words (at most one per link).
void ipc_primary_wait_many(dp_context* ctx, const std::vector<std::pair<int, size_t>>& pieces, cudaStream_t exec);
void ipc_send_rank(dp_context* ctx, dp_model* m, const dp_plan* plan, int primary, dp_run_stats* stats);
void ipc_close(dp_context* ctx);
void ipc_close_model(dp_model* m);
// The model's HBM slots on dev (infer.cu).
void acquire_slots(dp_context* ctx, dp_model* m, int dev, const int8_t* method);

}  // namespace dp
